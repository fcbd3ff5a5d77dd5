"""Write profiles/ncu_traffic_<workload>_<pattern>.json (read by bench.py's roofline block) from an
ncu --set full report of one counting launch: python tools/ncu_traffic.py REPORT.ncu-rep c5 k6_minus_e"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rep, workload, pattern = sys.argv[1:4]
prefix = os.path.join(ROOT, "profiles", f"r02_ncu_{workload}_{pattern}_final")
subprocess.check_call([sys.executable, os.path.join(ROOT, "tools", "ncu_summary.py"), rep, prefix],
                      stdout=subprocess.DEVNULL)
d = json.load(open(prefix + ".json"))


def val(k):
    return float(d[k]["value"].replace(",", ""))


unit = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
rate = {"byte/s": 1e-9, "Kbyte/s": 1e-6, "Mbyte/s": 1e-3, "Gbyte/s": 1.0, "Tbyte/s": 1e3}
out = {
    "workload": workload, "pattern": pattern,
    "kernel": f"stm_count_kernel (registers {d['launch__registers_per_thread']['value']}, grid "
              f"{d['launch__grid_size']['value']} x {d['launch__block_size']['value']})",
    "dram_bytes_per_launch": d["dram_bytes_per_launch"],
    "dram__bytes_read.sum": d["dram__bytes_read.sum"], "dram__bytes_write.sum": d["dram__bytes_write.sum"],
    "kernel_ms": val("gpu__time_duration.sum"),
    "warp_execution_efficiency": val("smsp__thread_inst_executed_per_inst_executed.ratio") / 32.0,
    "dram_read_gbs": val("dram__bytes_read.sum.per_second") * rate[d["dram__bytes_read.sum.per_second"]["unit"]],
    "l2_gbs": (val("lts__t_bytes.sum.per_second") * rate[d["lts__t_bytes.sum.per_second"]["unit"]]
               if "lts__t_bytes.sum.per_second" in d else val("lts__t_sectors.sum.per_second") * 32.0),  # sector/ns * 32 B
    "l2_hit_pct": val("lts__t_sector_hit_rate.pct"), "l1_hit_pct": val("l1tex__t_sector_hit_rate.pct"),
    "warps_active_pct": val("sm__warps_active.avg.pct_of_peak_sustained_active"),
    "top_stalls_per_issue": d["stalls_per_issue"],
    "source": f"ncu --set full --clock-control none --import-source on -k regex:stm_count_kernel -s 1 -c 1 "
              f"python tools/prof_run.py {workload} {pattern} (2nd launch); full summary {os.path.relpath(prefix, ROOT)}.json",
}
json.dump(out, open(os.path.join(ROOT, "profiles", f"ncu_traffic_{workload}_{pattern}.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
