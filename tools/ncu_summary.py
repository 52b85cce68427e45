#!/usr/bin/env python
"""Summarise one `ncu --set full` capture (one launch) into a committed JSON under profiles/.

Usage: python tools/ncu_summary.py REPORT.ncu-rep OUT.json --images N [--n-exc 6400] [--source TEXT]
bench.py reads profiles/ncu_full_latest.json for roofline.traffic when the launch shape matches."""
import argparse
import csv
import io
import json
import subprocess

KEYS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "lts__t_bytes.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.per_cycle_active", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "smsp__cycles_active.avg",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("out")
    ap.add_argument("--images", type=int, required=True)
    ap.add_argument("--n-exc", type=int, default=6400)
    ap.add_argument("--source", default="")
    a = ap.parse_args()
    txt = subprocess.run(["ncu", "-i", a.report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = dict(zip(hdr, vals))
    u = dict(zip(hdr, units))
    metrics = {k: [d[k], u[k]] for k in KEYS if k in d}

    def nbytes(k):
        return float(d[k].replace(",", "")) * SCALE.get(u[k], 1)
    out = {"kernel": d.get("Kernel Name", "?"), "images_per_launch": a.images, "n_exc": a.n_exc,
           "source": a.source or a.report,
           "dram_bytes_per_launch": nbytes("dram__bytes_read.sum") + nbytes("dram__bytes_write.sum"),
           "metrics": metrics}
    json.dump(out, open(a.out, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
