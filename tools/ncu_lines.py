"""Top source lines (and enclosing functions) of an ncu report by warp-stall samples.

python tools/ncu_lines.py report.ncu-rep [N] [--src-root DIR]
Reads the cuda,sass source page (needs -lineinfo builds and --import-source on); per line:
samples %, the three largest stall reasons, file:line, source. Then the same per function
(line ranges of the .cuh/.cu files found under --src-root, default the package csrc/)."""
import csv
import io
import os
import re
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def lines(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows, fname, header = [], None, None
    for rec in csv.reader(io.StringIO(out)):
        if not rec:
            continue
        if rec[0] == "File Path":
            fname = rec[1].split("/")[-1]
            continue
        if rec[0] == "Line No":
            header = rec
            continue
        if header is None or not rec[0].isdigit():
            continue
        try:
            smp = int(rec[4] or 0)
        except ValueError:
            continue
        stalls = {}
        for k, v in zip(header, rec):
            if k.startswith("stall_") and "Not Issued" not in k:
                try:
                    stalls[k[6:]] = int(v or 0)
                except ValueError:
                    pass
        rows.append((smp, fname, int(rec[0]), rec[1].strip(), stalls))
    return rows


def functions(src_root):
    """file -> sorted [(first line, function name)]"""
    fmap = {}
    pat = re.compile(r"^(?:template <[^>]*>\s*)?(?:__global__|__device__)[^(]*?\b(\w+)\s*\(")
    for dp, _, fs in os.walk(src_root):
        for f in fs:
            if not f.endswith((".cuh", ".cu")):
                continue
            starts = []
            for i, line in enumerate(open(os.path.join(dp, f)), 1):
                m = pat.match(line)
                if m:
                    starts.append((i, m.group(1)))
            fmap[f] = starts
    return fmap


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    src_root = os.path.join(ROOT, "paper_conf_icppw_zhangczsdhay23_b200", "csrc")
    if "--src-root" in sys.argv:
        src_root = sys.argv[sys.argv.index("--src-root") + 1]
    rows = lines(args[0])
    top = int(args[1]) if len(args) > 1 else 40
    tot = sum(r[0] for r in rows) or 1
    print(f"total stall samples {tot}")
    for smp, f, ln, src, st in sorted(rows, key=lambda r: -r[0])[:top]:
        reasons = " ".join(f"{k}:{100 * v / max(smp, 1):.0f}%" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:3] if v)
        print(f"{100 * smp / tot:5.1f}%  {f}:{ln:<5d} {src[:80]:80s} [{reasons}]")
    fmap = functions(src_root)
    agg = defaultdict(int)
    for smp, f, ln, _, _ in rows:
        name = "?"
        for start, fn in fmap.get(f, []):
            if start <= ln:
                name = fn
        agg[(f, name)] += smp
    print("\nper function (enclosing definition in the source; inlined code counts where it is written):")
    for (f, name), smp in sorted(agg.items(), key=lambda kv: -kv[1])[:25]:
        print(f"{100 * smp / tot:5.1f}%  {f}:{name}")


if __name__ == "__main__":
    main()
