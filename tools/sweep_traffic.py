"""Sum the DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of the
sweep-body kernels of one ncu launch list (tools/prof_sweep.py --what sweep1)
and write profiles/sweep_traffic.json, which bench.py reports as
roofline.traffic.  Binning kernels (classify, radix sort, plans) are excluded:
they run once per level, not per sweep.

    python tools/sweep_traffic.py profiles/r01_sweep1_c5_launches_v3.csv
"""
import csv
import json
import os
import sys

SWEEP = ("sweep_", "k_stage", "k_commit", "hub_coop", "k_part_", "k_tile_starts")


def main():
    path = sys.argv[1]
    data, order = {}, []
    hdr = None
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr):
            continue
        d = dict(zip(hdr, r))
        key = (int(d["ID"]), d["Kernel Name"])
        if key not in data:
            data[key] = {}
            order.append(key)
        data[key][d["Metric Name"]] = float(d["Metric Value"])
    tot, t_ms, nk = 0.0, 0.0, 0
    for k in order:
        name = k[1].replace("void ", "")
        if any(s in name for s in SWEEP):
            m = data[k]
            tot += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
            t_ms += m.get("gpu__time_duration.sum", 0) / 1e6
            nk += 1
    out = {"dram_bytes_per_sweep": tot, "kernels": nk, "ncu_time_ms": t_ms,
           "source": f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none "
                     f"(tools/prof_sweep.py --what sweep1), {os.path.basename(path)}"}
    dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "sweep_traffic.json")
    json.dump(out, open(dst, "w"), indent=1)
    print(out)


if __name__ == "__main__":
    main()
