"""Summarise .ncu-rep captures into profiles/ (text + JSON the bench reads for `roofline.traffic`).

usage: python scripts/ncu_summary.py <round tag> <key>[@<launch index>,...]=<report.ncu-rep> ...
  every launch of the report goes into profiles/ncu_<tag>.md; the traffic entry <key> (profiles/ncu_traffic.json,
  read by bench.py) takes the launch given after '@' (default: the last one), or several as key1@i,key2@j
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__bytes_read.sum.per_second", "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum",
        "syslts__t_sector_hit_rate.pct", "pcie__read_bytes.sum.per_second", "pcie__write_bytes.sum.per_second",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warp_latency_per_inst_issued.ratio", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__occupancy_limit_registers", "sm__maximum_warps_per_active_cycle_pct",
        "smsp__inst_executed.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3,
         "msecond": 1e-3, "s": 1}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, vals):
            d[h] = (v, u)
        res.append(d)
    return res


def num(d, key):
    if key not in d:
        return None
    v, u = d[key]
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return None
    return x * SCALE.get(u, 1)


def main():
    tag = sys.argv[1]
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    md = [f"# ncu summary — {tag}", ""]
    for arg in sys.argv[2:]:
        if arg.startswith("--"):
            continue
        q, rep = arg.split("=", 1)
        picks = {}  # launch index -> traffic key
        for part in q.split(","):
            key, _, idx = part.partition("@")
            picks[int(idx) if idx else -1] = key
        launches = raw(rep)
        if -1 in picks:
            picks[len(launches) - 1] = picks.pop(-1)
        for i, d in enumerate(launches):
            name = d.get("Kernel Name", ("?", ""))[0]
            dur = num(d, "gpu__time_duration.sum")
            rd, wr = num(d, "dram__bytes_read.sum"), num(d, "dram__bytes_write.sum")
            sysr = num(d, "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum")
            md.append(f"## {picks.get(i, q)}: `{name}` (launch {i})")
            md.append("")
            md.append("| metric | value | unit |")
            md.append("|---|---|---|")
            for k in KEYS:
                if k in d:
                    md.append(f"| {k} | {d[k][0]} | {d[k][1]} |")
            if dur:
                md.append("")
                md.append(f"derived: DRAM traffic {((rd or 0) + (wr or 0)) / 1e6:.1f} MB/launch, "
                          f"{((rd or 0) + (wr or 0)) / dur / 1e9:.1f} GB/s; sysmem (zero-copy) reads "
                          f"{(sysr or 0) * 32 / 1e9:.3f} GB/launch = {(sysr or 0) * 32 / dur / 1e9:.1f} GB/s")
            md.append("")
            if i in picks:
                traffic[picks[i]] = {"kernel": name, "dram_bytes": (rd or 0) + (wr or 0),
                                     "sysmem_read_bytes": (sysr or 0) * 32, "duration_s": dur, "tag": tag}
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"ncu_{tag}.md"), "w") as f:
        f.write("\n".join(md) + "\n")
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
