"""Summarise an ncu --set full report (raw page + top source lines) into JSON/text for profiles/.

usage: python tools/ncu_summary.py REPORT.ncu-rep OUT_PREFIX
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "l1tex__t_bytes.sum", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__inst_executed.avg.per_cycle_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum.per_second",
        "l1tex__t_bytes.sum.per_second", "dram__bytes_read.sum.per_second", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "lts__t_sectors.sum",
        "lts__t_sectors.sum.per_second"]


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u, v = rows[0], rows[1], rows[2]
    res = {}
    stalls = {}
    for i, name in enumerate(h):
        if name in KEYS:
            res[name] = {"unit": u[i], "value": v[i]}
        if name.startswith("smsp__average_warps_issue_stalled_") and name.endswith("_per_issue_active.ratio"):
            try:
                stalls[name[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]] = float(v[i])
            except ValueError:
                pass
    res["stalls_per_issue"] = dict(sorted(stalls.items(), key=lambda x: -x[1])[:10])

    def num(k, scale):
        x = res[k]
        f = float(x["value"].replace(",", ""))
        return f * scale.get(x["unit"], 1.0)
    sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    res["dram_bytes_per_launch"] = num("dram__bytes_read.sum", sc) + num("dram__bytes_write.sum", sc)
    res["report"] = rep
    json.dump(res, open(out + ".json", "w"), indent=1)
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    iS = hdr.index("Warp Stall Sampling (All Samples)")
    lines = []
    for r in rows:
        if len(r) > iS and r[0] not in ("", "Line No"):
            try:
                lines.append((int(r[iS]), int(r[0]), r[1].strip()[:110]))
            except ValueError:
                pass
    lines.sort(reverse=True)
    tot = sum(x[0] for x in lines) or 1
    with open(out + "_hot_lines.txt", "w") as f:
        f.write(f"# warp-stall samples per kernel.cu line (top 40 of {tot}) from {rep}\n")
        for s, ln, t in lines[:40]:
            f.write(f"{s:8d} {100.0 * s / tot:5.1f}%  kernel.cu:{ln:<5d} {t}\n")
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
