#!/usr/bin/env python
"""Per-stage instruction shares of the step kernel (the Fig. 13(c) analogue
for the optimised kernel, PAPER.md L406-L408 / L496-L504): every executed
SASS instruction of an `ncu --set full` capture is attributed to the
innermost source line it was compiled from (nvdisasm -gi line info of the
same libsharp.so), and that line to a stage of the method by its text.

usage: tools/stage_shares.py REPORT.ncu-rep PIXELS OUT.json [KERNEL_SUBSTR]
Writes {"kernel", "thread_instr_per_px", "shares": {stage: {"thread_instr_per_px", "share"}},
"source_sha256"} and prints a table."""
import collections
import csv
import glob
import importlib.util
import io
import json
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..")
CSRC = os.path.join(ROOT, "paper_conf_icpp_fanjzac15_b200", "csrc")

# (stage, keywords of the source line) -- first match wins
RULES = [
    ("table build (strength / oscStrength, L178 L184)", ["lut_entry", "lut_adj", "lut_osc", "frame_mean", "pow(", "exp("]),
    ("pass-1 accumulation + reduction (L174)", ["fma_f32_f16", "__reduce_add_sync", "atomicAdd(&sp.acc", "sum = __fadd_rn",
                                                "vmask", "acc[x]", "acc[i]", "sum += acc",
                                                "r >= 1 && r + 2 <= rmax1"]),
    ("Sobel (L158-L172)", ["hsub(", "hfma(kTwo", "habsadd", "sobel(", "gx =", "gy =", "add.u32", "d.s[i]"]),
    ("3x3 max / min (L182)", ["__vimax3", "__vimin3"]),
    ("unpack + neighbour exchange", ["kMinus1024", "kF16Bias", "__shfl_sync(0xffffffffu, O1", "__shfl_sync(0xffffffffu, E0",
                                    "prmt(PO", "prmt(O0", "prmt(E0", "prmt(E1", "row_words", "lds_u64"]),
    ("downscale (L130)", ["dblock", "blk4", "__dp4a", "dm1", "d2 ="]),
    ("upscale body (L146)", ["lin2", "cwt(", "f4fma", "f4add", "f4twice_diff", "slope", "mul.rn.f32x2", "fma.rn.f32x2",
                            "f2pack", "f2unpack", "NU[8]", "nu01", "nu23", "nu45", "nu67"]),
    ("upscale border + frame (L140-L142, L160, L208)", ["ring_rows", "ring_cols", "set_frame_px", "line_val", "div16",
                                                        "set_px", "u[", "NU[x] = -u"]),
    ("strength lookup (L178)", ["q8", "lds_f2", "lut_q"]),
    ("pError + preliminary (L148, L178)", ["rb.c[p]", "__fmaf_rn(L.x", "P[x] ="]),
    ("overshoot (L180-L212)", ["fminf(fmaxf", "mxf", "mnf", "sub2", "__fmaf_rn(osc", "T8[x]", "add.rn.f32x2",
                               "sub.rn.f32x2"]),
    ("output (R14)", ["pack4_rni_u8", "cvt.", "st_stream", "orow", "uint2 o"]),
]
PIPE = "pipeline (TMA, barriers, scheduling, loop control)"


def classify(text):
    for stage, keys in RULES:
        if any(k in text for k in keys):
            return stage
    return PIPE


def main():
    rep, px, out = sys.argv[1], float(sys.argv[2]), sys.argv[3]
    fsub = sys.argv[4] if len(sys.argv) > 4 else "step_kernelILb0"
    lib = os.path.join(ROOT, "paper_conf_icpp_fanjzac15_b200", "libsharp.so")
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=tmp, check=True, capture_output=True)
    sass = ""
    for cub in glob.glob(os.path.join(tmp, "*.cubin")):
        t = subprocess.run(["nvdisasm", "-gi", "-c", cub], capture_output=True, text=True).stdout
        if fsub in t:
            sass = t
            break
    if not sass:
        sys.exit(f"{fsub} not found in {lib}")
    # address -> innermost (file, line)
    # (a group of //## lines precedes an instruction; its FIRST line is the
    # innermost inlined location)
    # The whole inline chain is kept: classification walks from the innermost
    # frame outwards to the first line a rule recognises (intrinsic headers and
    # one-line helpers such as hadd() match no rule and are skipped).
    attr, infunc, chain, fresh = {}, False, [], True
    for line in sass.splitlines():
        if line.startswith(".text.") or "//----" in line:
            infunc = fsub in line
        if not infunc:
            continue
        m = re.match(r'\s*//## File "([^"]+)", line (\d+)', line)
        if m:
            if fresh:
                chain = []
                fresh = False
            chain.append((m.group(1).split("/")[-1], int(m.group(2))))
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
        if m:
            fresh = True
            if chain:
                attr[int(m.group(1), 16)] = tuple(chain)
    # executed warp-instructions per address
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hdr = rows[1]
    ia, iex = hdr.index("Address"), hdr.index("Instructions Executed")
    recs = [(int(r[ia], 16), int(r[iex] or 0)) for r in rows[2:] if len(r) > iex]
    base = recs[0][0]
    files = {}

    def text(f, ln):
        if f not in files:
            p = os.path.join(CSRC, f)
            files[f] = open(p).read().splitlines() if os.path.exists(p) else []
        L = files[f]
        return L[ln - 1] if 0 < ln <= len(L) else f
    def stage_of(chain):
        for f, ln in chain:
            if not os.path.exists(os.path.join(CSRC, f)):
                if "math" in f or "libdevice" in f:  # libm pow / exp: the table build
                    return RULES[0][0]
                continue
            for stage, keys in RULES:
                if any(k in text(f, ln) for k in keys):
                    return stage
        return PIPE
    by = collections.Counter()
    for a, e in recs:
        ch = attr.get(a - base)
        by[stage_of(ch) if ch else PIPE] += e
    tot = sum(by.values())
    shares = {k: {"thread_instr_per_px": 32 * v / px, "share": v / tot} for k, v in by.most_common()}
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    bench = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bench)
    res = {"kernel": fsub, "report": os.path.basename(rep), "pixels": px, "thread_instr_per_px": 32 * tot / px,
           "shares": shares, "kernel_kind": "step", "source_sha256": bench.kernel_source_hash("step"),
           "method": "ncu Instructions Executed per SASS address, attributed by nvdisasm -gi to the innermost "
                     "source line, classified by the line's text (tools/stage_shares.py RULES)"}
    json.dump(res, open(out, "w"), indent=1)
    print(f"{32 * tot / px:.2f} thread-instr/px")
    for k, v in shares.items():
        print(f"  {k:52s} {v['thread_instr_per_px']:6.2f}/px  {v['share']:6.1%}")


if __name__ == "__main__":
    main()
