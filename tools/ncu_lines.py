"""Top source lines of an ncu report by warp-stall samples (cuda,sass source page).

python tools/ncu_lines.py report.ncu-rep [N]   -> samples %, file:line, source"""
import csv
import io
import subprocess
import sys


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
        rows.append((smp, fname, int(rec[0]), rec[1].strip()))
    return rows


def main():
    rows = lines(sys.argv[1])
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    tot = sum(r[0] for r in rows) or 1
    print(f"total stall samples {tot}")
    for smp, f, ln, src in sorted(rows, reverse=True)[:top]:
        print(f"{100 * smp / tot:5.1f}%  {f}:{ln:<5d} {src[:110]}")


if __name__ == "__main__":
    main()
