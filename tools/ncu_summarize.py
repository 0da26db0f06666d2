"""Summarise ncu captures into profiles/ (run here, on the CPU box).

python tools/ncu_summarize.py <rep.ncu-rep | raw.csv> <workload key> <alg_bytes_per_launch> [out_dir]

Appends/updates profiles/ncu_summary.json[key] with the per-launch DRAM bytes,
duration and throughput of the captured band-kernel launch(es), and writes a
text dump of the key metrics next to it.
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__average_warp_latency_per_inst_issued.ratio", "launch__shared_mem_per_block_dynamic"]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
        "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "nsecond": 1e-9}


def main():
    rep, key, alg = sys.argv[1], sys.argv[2], float(sys.argv[3])
    out_dir = sys.argv[4] if len(sys.argv) > 4 else "profiles"
    if rep.endswith(".csv"):          # `ncu -i X --page raw --csv` exported on the GPU box
        raw = open(rep).read()
    else:
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                             text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        if "sat_band_kernel" not in d.get("Kernel Name", ""):
            continue
        m = {}
        for k in KEYS:
            if k in d:
                u = units[hdr.index(k)]
                v = float(d[k].replace(",", ""))
                m[k] = v * UNIT.get(u, 1.0)
        launches.append(m)
    if not launches:
        sys.exit("no sat_band_kernel launch in " + rep)
    n = len(launches)
    avg = {k: sum(l.get(k, 0.0) for l in launches) / n for k in KEYS}
    dram = avg["dram__bytes_read.sum"] + avg["dram__bytes_write.sum"]
    t = avg["gpu__time_duration.sum"]
    entry = {"report": os.path.basename(rep), "launches": n,
             "dram_bytes_per_launch": dram,
             "dram_read_bytes": avg["dram__bytes_read.sum"],
             "dram_write_bytes": avg["dram__bytes_write.sum"],
             "alg_bytes_per_launch": alg, "traffic_over_alg": dram / alg,
             "duration_s_under_ncu": t, "dram_gbs_under_ncu": dram / t / 1e9,
             "dram_pct_peak": avg["dram__throughput.avg.pct_of_peak_sustained_elapsed"],
             "registers": avg["launch__registers_per_thread"], "grid": avg["launch__grid_size"],
             "block": avg["launch__block_size"],
             "smem_dyn": avg.get("launch__shared_mem_per_block_dynamic")}
    os.makedirs(out_dir, exist_ok=True)
    p = os.path.join(out_dir, "ncu_summary.json")
    allj = json.load(open(p)) if os.path.exists(p) else {}
    allj[key] = entry
    json.dump(allj, open(p, "w"), indent=1, sort_keys=True)
    print(json.dumps({key: entry}, indent=1))


if __name__ == "__main__":
    main()
