#!/usr/bin/env python
"""Per-CUDA-source-line warp-stall attribution from an ncu report captured with --import-source on
(and -lineinfo).  Usage: python tools/ncu_lines.py report.ncu-rep [top_n]"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 50
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    cur, hdr, recs = None, None, []
    for r in csv.reader(io.StringIO(txt)):
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr and r[0].isdigit():
            try:
                recs.append((cur, int(r[0]), r[1], float(r[4] or 0), float(r[5] or 0), float(r[7] or 0)))
            except (ValueError, IndexError):
                pass
    tot = sum(x[3] for x in recs) or 1.0
    print(f"total stall samples {tot:.0f}")
    for f, ln, src, s_all, s_ni, inst in sorted(recs, key=lambda x: -x[3])[:top]:
        print(f"{100 * s_all / tot:5.1f}%  (not-issued {100 * s_ni / tot:4.1f}%)  inst {inst:>10.0f}  {f[:16]}:{ln:<5} {src.strip()[:90]}")


if __name__ == "__main__":
    main()
