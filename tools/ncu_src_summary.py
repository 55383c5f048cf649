"""Per-source-line warp-stall summary of an `ncu --set full --import-source on` capture.

    python tools/ncu_src_summary.py <kernel substring> <report.ncu-rep> [lines] > summary.md

Maps the SASS offsets of the report's source page to CUDA source lines with the line table
of the in-tree libpsim.so (nvdisasm --print-line-info; the .so must be the build that was
profiled; PSIM_LIB / PSIM_CSRC point at another build and its sources) and prints the lines with
the most stall samples and their top stall reasons."""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.environ.get("PSIM_CSRC") or os.path.join(ROOT, "paper_conf_sc_pandeylfhl22_b200", "csrc")


def line_table(kern):
    lib = os.environ.get("PSIM_LIB") or os.path.join(ROOT, "paper_conf_sc_pandeylfhl22_b200", "libpsim.so")
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=d, capture_output=True, check=True)
        sass = ""
        for f in sorted(os.listdir(d)):
            if f.endswith(".cubin"):
                sass += subprocess.run(["nvdisasm", "--print-line-info", os.path.join(d, f)],
                                       capture_output=True, text=True).stdout
    lines = sass.split("\n")
    start = [i for i, l in enumerate(lines) if l.startswith(".text._ZN4psim") and kern in l][0]
    off2line, cur = {}, None
    for l in lines[start + 1:]:
        if l.startswith(".text.") or l.startswith("//---") or l.lstrip().startswith(".section"):
            break                                   # next function / section / cubin
        m = re.search(r'//## File "([^"]+)", line (\d+)', l)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.search(r"/\*([0-9a-f]{4,})\*/", l)
        if m and cur:
            off2line[int(m.group(1), 16)] = cur
    return off2line


def main():
    kern, rep = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    idx = {h: i for i, h in enumerate(hdr)}
    data = [r for r in rows[2:] if len(r) >= len(hdr)]
    base = int(data[0][0], 16)
    off2line = line_table(kern)
    stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    agg = collections.defaultdict(collections.Counter)
    tot = 0
    for r in data:
        ln = off2line.get(int(r[0], 16) - base, ("?", 0))
        s = int(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
        tot += s
        agg[ln]["samples"] += s
        agg[ln]["inst"] += int(r[idx["Instructions Executed"]] or 0)
        for c in stall_cols:
            v = int(r[idx[c]] or 0)
            if v:
                agg[ln][c] += v
    src = {}
    for f in os.listdir(CSRC):
        src[f] = open(os.path.join(CSRC, f)).read().split("\n")
    print(f"# ncu source-level stall summary: `{kern}` ({os.path.basename(rep)})\n")
    print(f"Total warp-stall samples: {tot}.  Columns: samples, warp instructions executed, source line, "
          f"top stall reasons.\n")
    print("| samples | share | instructions | line | source | top stalls |\n|---|---|---|---|---|---|")
    for ln, c in sorted(agg.items(), key=lambda x: -x[1]["samples"])[:top]:
        st = sorted(((v, k) for k, v in c.items() if k not in ("samples", "inst")), reverse=True)[:3]
        f = src.get(ln[0])
        text = f[ln[1] - 1].strip()[:70].replace("|", "\\|") if f and 0 < ln[1] <= len(f) else ""
        print(f"| {c['samples']} | {100 * c['samples'] / max(tot, 1):.1f}% | {c['inst']} | {ln[0]}:{ln[1]} | `{text}` | "
              + ", ".join(f"{k.replace('stall_', '')} {v}" for v, k in st) + " |")


if __name__ == "__main__":
    main()
