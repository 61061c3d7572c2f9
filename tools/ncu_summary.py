"""Summarise an ncu report (read here, no GPU needed) into profiles/.

    python tools/ncu_summary.py gpurun_out/prof_c2.ncu-rep profiles/r1_ncu_c2

Writes <out>.json (per launch: kernel, duration, DRAM bytes read/written,
throughput percentages, occupancy, registers, top stall reasons) and
<out>.md (a table).  Also merges the per-kernel mean DRAM bytes per launch into
profiles/ncu_traffic.json, which bench.py reports as roofline.traffic.
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration_us",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "dram__bytes.sum.per_second": "dram_bytes_per_s",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "launch__shared_mem_per_block_dynamic": "dyn_smem",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "fma_pipe_pct",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active": "xu_pipe_pct",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active": "tensor_pipe_pct",
    "lts__t_sectors_op_atom.sum": "l2_atom_sectors",
    "smsp__inst_executed.sum": "inst_executed",
}
def _hbm_gbs():
    for p in ("MEASURED_PEAKS.json", os.path.join(os.path.dirname(__file__), "..", "MEASURED_PEAKS.json")):
        if os.path.exists(p):
            return float(json.load(open(p))["hbm_gbs"])
    return 6465.8   # the driver's measured figure on this pool (MEASURED_PEAKS.json, round 1)


HBM_GBS = _hbm_gbs()
B = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}
UNIT = {"dram_read": B, "dram_write": B,
        "duration_us": {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "ns": 1e-3, "us": 1.0, "ms": 1e3}}


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    head, units = rows[0], rows[1]
    stall_cols = [i for i, h in enumerate(head) if h.startswith("smsp__average_warps_issue_stalled_")
                  and h.endswith("_per_issue_active.ratio")]
    launches = []
    for r in rows[2:]:
        d = {"kernel": r[head.index("Kernel Name")]}
        for k, name in KEYS.items():
            if k in head:
                i = head.index(k)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                v *= UNIT.get(name, {}).get(units[i], 1.0)
                d[name] = v
        if "dram_pct" not in d and d.get("duration_us"):
            # no throughput metric in the capture: DRAM bytes / duration against the measured peak
            d["dram_pct"] = 100.0 * (d.get("dram_read", 0) + d.get("dram_write", 0)) / (d["duration_us"] * 1e-6) / (HBM_GBS * 1e9)
        stalls = []
        for i in stall_cols:
            try:
                stalls.append((float(r[i].replace(",", "")), head[i]))
            except ValueError:
                pass
        stalls.sort(reverse=True)
        d["top_stalls"] = [[h.split("stalled_")[-1].replace("_per_issue_active.ratio", ""), round(v, 2)]
                           for v, h in stalls[:5]]
        launches.append(d)
    write(launches, os.path.basename(rep), out)


def write(launches, rep_name, out):
    for d in launches:
        if d.get("dram_pct") is None and d.get("duration_us"):
            d["dram_pct"] = 100.0 * (d.get("dram_read", 0) + d.get("dram_write", 0)) / (d["duration_us"] * 1e-6) / (HBM_GBS * 1e9)
    json.dump({"report": rep_name, "launches": launches}, open(out + ".json", "w"), indent=1)
    rep = rep_name
    with open(out + ".md", "w") as f:
        f.write("# ncu summary: %s\n\n" % os.path.basename(rep))
        f.write("| kernel | us | DRAM read MB | DRAM write MB | DRAM % | SM % | occ % | regs | grid | top stalls |\n")
        f.write("|---|---|---|---|---|---|---|---|---|---|\n")
        for d in launches:
            f.write("| %s | %.1f | %.1f | %.1f | %.1f | %.1f | %.1f | %d | %d | %s |\n" % (
                d["kernel"][:60], d.get("duration_us", 0), d.get("dram_read", 0) / 1e6, d.get("dram_write", 0) / 1e6,
                d.get("dram_pct", 0), d.get("sm_pct", 0), d.get("achieved_occupancy_pct", 0), d.get("regs", 0),
                d.get("grid", 0), ", ".join("%s %.1f" % (a, b) for a, b in d["top_stalls"][:3])))
    traffic_path = os.path.join(os.path.dirname(out) or ".", "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    per = {}
    for d in launches:
        nm = d["kernel"].replace("void ", "").split("(")[0].replace("slate::", "")
        nm = nm.replace("<slate::", "<")
        per.setdefault(nm, []).append(d.get("dram_read", 0) + d.get("dram_write", 0))
    for nm, v in per.items():
        traffic[nm] = sum(v) / len(v)
    json.dump(traffic, open(traffic_path, "w"), indent=1)
    print(open(out + ".md").read())


if __name__ == "__main__":
    if sys.argv[1] == "--from-json":   # re-render a summary already extracted (the .ncu-rep is scratch)
        j = json.load(open(sys.argv[2] + ".json"))
        write(j["launches"], j["report"], sys.argv[2])
    else:
        main(sys.argv[1], sys.argv[2])
