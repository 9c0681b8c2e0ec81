#!/usr/bin/env python
"""Summarise ncu reports (.ncu-rep) and launch lists into profiles/ (text + JSON, committed).

  python scripts/ncu_summary.py --tag r01 --config lofar gpurun_out/prof_gridder_X.ncu-rep ... \
         [--launches gpurun_out/launches_X.csv]
"""
import argparse
import csv
import io
import json
import os
import re
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "sm clock"),
    ("launch__grid_size", "grid"), ("launch__block_size", "block"),
    ("launch__registers_per_thread", "registers/thread"),
    ("sm__warps_active.avg.per_cycle_active", "active warps/SM"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU (MUFU) pipe %"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("dram__bytes_read.sum", "DRAM read"), ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_bytes.sum", "L2 bytes"),
]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return [dict(zip(rows[0], zip(rows[1], r))) for r in rows[2:]]


def summarize(rep):
    res = []
    for d in raw(rep):
        name = d.get("Kernel Name", ("", "?"))[1]
        rec = {"kernel": name}
        for k, label in KEYS:
            if k in d:
                u, v = d[k]
                rec[label] = f"{v} {u}".strip()
        st = []
        for h, (u, v) in d.items():
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    st.append((float(v), h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        rec["top stalls (per issue)"] = ", ".join(f"{n} {v:.2f}" for v, n in sorted(st, reverse=True)[:6])
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            if k in d:
                u, v = d[k]
                b += float(v.replace(",", "")) * SCALE.get(u, 1)
        rec["dram_bytes"] = b
        # per-pipe utilisation: instructions issued to a pipe and cycles the pipe was busy, both as % of its
        # peak (ComputeWorkloadAnalysis); the binding pipe is the busiest of them
        pipes = {}
        for h, (u, v) in d.items():
            m = re.match(r"^sm__(inst_executed_pipe|pipe)_([a-z0-9_]+?)(_cycles_active)?"
                         r"\.avg\.pct_of_peak_sustained_active$", h)
            if not m:
                continue
            try:
                val = float(v.replace(",", ""))
            except ValueError:
                continue
            key = ("inst:" if m.group(1) == "inst_executed_pipe" else "cycles:") + m.group(2)
            pipes[key] = val
        if pipes:
            rec["pipes %"] = ", ".join(f"{k} {v:.1f}" for k, v in sorted(pipes.items(), key=lambda x: -x[1])[:12])
            bk = max(pipes, key=pipes.get)
            rec["binding pipe"] = f"{bk} {pipes[bk]:.1f}%"
            rec["_pipes"] = pipes
        ph = loop_share(rep, name)
        if ph is not None:
            rec["inner-loop share of stall samples"] = f"{100 * ph:.1f}% (per-item prologue / epilogue: {100 * (1 - ph):.1f}%)"
            rec["_loop_share"] = ph
        ia = d.get("smsp__issue_active.avg.pct_of_peak_sustained_active")
        if ia:
            rec["_issue"] = float(ia[1].replace(",", ""))
        res.append(rec)
    return res


def loop_share(rep, kernel_name):
    """Share of the warp-stall samples in the kernel's inner loop: SASS instructions executed at least 5% as
    often as the most executed one (per-item code -- setup, A-term / taper, subgrid DFT, adder / splitter,
    stores -- runs ~100x less often).  None without a source page."""
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    try:
        hi = next(i for i, r in enumerate(rows) if "# Samples" in r and "Instructions Executed" in r)
    except StopIteration:
        return None
    hdr = rows[hi]
    si, ei = hdr.index("# Samples"), hdr.index("Instructions Executed")
    data = []
    for r in rows[hi + 1:]:
        if len(r) <= max(si, ei):
            continue
        try:
            data.append((float(r[si]), float(r[ei])))
        except ValueError:
            continue
    if not data:
        return None
    mx = max(e for _, e in data)
    tot = sum(smp for smp, _ in data)
    return sum(smp for smp, e in data if e >= 0.05 * mx) / tot if tot else None


def launches(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    idx = {h: i for i, h in enumerate(hdr)}
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[start + 1:]:
        if len(r) < len(hdr) or r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        v = float(r[idx["Metric Value"]].replace(",", ""))
        v *= {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}.get(r[idx["Metric Unit"]], 1.0)
        k = r[idx["Kernel Name"]].split("(")[0][:70]
        agg[k][0] += 1
        agg[k][1] += v
    tot = sum(v[1] for v in agg.values())
    return [(k, n, ms, 100 * ms / tot) for k, (n, ms) in sorted(agg.items(), key=lambda x: -x[1][1])]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("reports", nargs="*")
    ap.add_argument("--tag", required=True)
    ap.add_argument("--config", default="lofar")
    ap.add_argument("--launches")
    ap.add_argument("--note", default="")
    ap.add_argument("--capture-timesteps", type=int, default=0,
                    help="T of the captured workload (bench.py scales dram_bytes to its own T)")
    ap.add_argument("--bench", help="bench.py JSON line of the same build: adds its CUDA-event shares")
    args = ap.parse_args()
    md = [f"# ncu summary {args.tag} ({args.config})", ""]
    if args.note:
        md += [args.note, ""]
    js_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    js = json.load(open(js_path)) if os.path.exists(js_path) else {}
    for rep in args.reports:
        for rec in summarize(rep):
            md.append(f"## {rec['kernel']}  ({os.path.basename(rep)})")
            for k, v in rec.items():
                if k != "kernel" and not k.startswith("_"):
                    md.append(f"- {k}: {v}")
            md.append("")
            short = "degridder" if "degridder" in rec["kernel"] else "gridder" if "gridder" in rec["kernel"] \
                else rec["kernel"].split("(")[0]
            ent = {"tag": args.tag, "kernel": rec["kernel"], "dram_bytes": rec["dram_bytes"]}
            if args.capture_timesteps:
                ent["capture_timesteps"] = args.capture_timesteps
            if "_pipes" in rec:
                p = rec["_pipes"]
                bk = max(p, key=p.get)
                ent.update({"binding_pipe": bk, "binding_pipe_frac": p[bk] / 100.0,
                            "inner_loop_sample_share": rec.get("_loop_share"),
                            "issue_active_frac": rec.get("_issue", 0.0) / 100.0,
                            "pipes_pct_of_peak": dict(sorted(p.items(), key=lambda x: -x[1]))})
            js.setdefault(args.config, {})[short] = ent
    if args.launches:
        md += ["## launch list (ncu gpu__time_duration, cold/serialised: compare shares)", "",
               "| kernel | launches | total ms | share |", "|---|---|---|---|"]
        rows = launches(args.launches)
        for k, n, ms, sh in rows:
            md.append(f"| `{k}` | {n} | {ms:.3f} | {sh:.1f}% |")
        # the timed step = grid zeroing + gridder + degridder; the rho benchmarks run after it
        step = [(k, n, ms) for k, n, ms, _ in rows if "gridder" in k or "FillFunctor" in k]
        tot = sum(ms / n for _, n, ms in step)
        bench = json.load(open(args.bench)).get("kernels", {}) if args.bench else {}
        md += ["", "Share of the timed step (fill + gridder + degridder), ncu launch list vs bench.py CUDA events:", "",
               "| kernel | mean ms / launch (ncu) | share (ncu) | share (bench) |", "|---|---|---|---|"]
        for k, n, ms in step:
            short = "degridder" if "degridder" in k else "gridder" if "gridder" in k else None
            b = bench.get(short, {}).get("share_of_step") if short else None
            md.append(f"| `{k}` | {ms / n:.3f} | {ms / n / tot:.4f} | {'-' if b is None else f'{b:.4f}'} |")
    open(os.path.join(ROOT, "profiles", f"{args.tag}_ncu_summary.md"), "w").write("\n".join(md) + "\n")
    json.dump(js, open(js_path, "w"), indent=1)


if __name__ == "__main__":
    main()
