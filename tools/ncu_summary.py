#!/usr/bin/env python
"""Summarise an ncu report (and optionally a launch-list CSV) into the
markdown / JSON files committed under profiles/<round>/.

usage: tools/ncu_summary.py REPORT.ncu-rep PIXELS_PER_LAUNCH OUT_DIR [LAUNCHES.csv]
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__inst_executed.sum",
    "sm__inst_executed.sum.per_cycle_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.avg.per_cycle_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "lts__t_sector_hit_rate.pct",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
]


def raw(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    recs = []
    for r in rows[2:]:
        d = {}
        for k in hdr:
            i = hdr.index(k)
            d[k] = (r[i], units[i])
        recs.append(d)
    return hdr, recs


def num(v):
    return float(v.replace(",", ""))


def main():
    report, px, out_dir = sys.argv[1], float(sys.argv[2]), sys.argv[3]
    os.makedirs(out_dir, exist_ok=True)
    hdr, recs = raw(report)
    stall_keys = [k for k in hdr if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")]
    lines = ["# ncu summary", "", f"report: `{os.path.basename(report)}`", ""]
    summary = []
    for rec in recs:
        name = rec.get("Kernel Name", ("?", ""))[0]
        lines += [f"## {name}", "", "| metric | value | unit |", "|---|---|---|"]
        for k in KEYS:
            if k in rec:
                lines.append(f"| {k} | {rec[k][0]} | {rec[k][1]} |")
        rd = num(rec["dram__bytes_read.sum"][0]) if "dram__bytes_read.sum" in rec else 0.0
        wr = num(rec["dram__bytes_write.sum"][0]) if "dram__bytes_write.sum" in rec else 0.0
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rd *= scale.get(rec["dram__bytes_read.sum"][1], 1)
        wr *= scale.get(rec["dram__bytes_write.sum"][1], 1)
        lines += ["", f"DRAM traffic per output pixel: {(rd + wr) / px:.3f} B "
                      f"(read {rd / px:.3f}, write {wr / px:.3f}; algorithmic 2.000)", ""]
        stalls = sorted(((num(rec[k][0]) if rec[k][0] else 0.0, k) for k in stall_keys), reverse=True)[:10]
        tot = sum(v for v, _ in stalls) or 1.0
        lines += ["warp-stall samples (top 10):", "", "| reason | samples | share |", "|---|---|---|"]
        for v, k in stalls:
            lines.append(f"| {k.replace('smsp__pcsamp_warps_issue_stalled_', '')} | {int(v)} | {v / tot:.1%} |")
        lines.append("")
        ent = {"kernel": name, "dram_read_bytes": rd, "dram_write_bytes": wr,
               "pixels_per_launch": px, "dram_bytes_per_px": (rd + wr) / px}
        # issue-rate evidence (the kernel is instruction-issue bound)
        for k, key in [("smsp__inst_executed.sum", "warp_instr"), ("gpu__time_duration.sum", "duration"),
                       ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active_pct"),
                       ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "fma_pipe_pct"),
                       ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "alu_pipe_pct")]:
            if k in rec and rec[k][0]:
                v = num(rec[k][0])
                if key == "warp_instr":
                    v *= {"inst": 1, "Kinst": 1e3, "Minst": 1e6, "Ginst": 1e9}.get(rec[k][1], 1)
                    ent["warp_instr_per_px"] = v / px
                    ent["thread_instr_per_px"] = 32 * v / px
                elif key == "duration":
                    v *= {"ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1}.get(rec[k][1], 1e-9)
                    ent["duration_s"] = v
                else:
                    ent[key] = v
        if "warp_instr_per_px" in ent:
            lines += [f"instructions: {ent['thread_instr_per_px']:.2f} thread-instr per output pixel "
                      f"({ent['warp_instr_per_px']:.4f} warp-instr/px)", ""]
        summary.append(ent)
    if len(sys.argv) > 4:
        lines += ["## launch list (ncu gpu__time_duration, cold-cache, serialised)", "", "```"]
        lines += open(sys.argv[4]).read().strip().splitlines()[-12:]
        lines += ["```", ""]
    open(os.path.join(out_dir, "ncu_summary.md"), "w").write("\n".join(lines))
    if summary:
        # keyed on the kernel's sources, so bench.py reports it only while they are unchanged
        sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
        import importlib.util
        spec = importlib.util.spec_from_file_location("bench", os.path.join(os.path.dirname(__file__), "..", "bench.py"))
        bench = importlib.util.module_from_spec(spec)
        spec.loader.exec_module(bench)
        kind = "res" if "res_kernel" in summary[0]["kernel"] else "step"
        summary[0]["kernel_kind"] = kind
        summary[0]["source_sha256"] = bench.kernel_source_hash(kind)
        name = "traffic.json" if kind == "step" else f"traffic_{kind}.json"
        json.dump(summary[0], open(os.path.join(out_dir, name), "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
