"""Summarise an `ncu --set full` report (exported with --page raw --csv): per kernel
launch the duration, DRAM bytes, PCIe bytes (rate x duration), sysmem sectors, occupancy
and the top stall reasons; also writes profiles/ncu_traffic.json (per kernel family, the
mean measured traffic per launch: DRAM bytes for HBM-bound kernels, PCIe bytes for the
host-link-bound gather/flush: the sysmem sectors, next to their DRAM bytes) which bench.py
reports as roofline.traffic / roofline.host_link_traffic."""
import collections
import csv
import json
import sys


def conv(v, unit):
    v = float(v) if v else 0.0
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
                "msecond": 1e-3, "ms": 1e-3, "nsecond": 1e-9, "Gbyte/s": 1e9, "Mbyte/s": 1e6, "Kbyte/s": 1e3,
                "byte/s": 1, "sector": 32}.get(unit, 1)


def main(raw_csv, out_txt, out_json):
    rows = list(csv.reader(open(raw_csv)))
    h, units, data = rows[0], rows[1], rows[2:]
    col = {n: i for i, n in enumerate(h)}
    stall = [i for i, x in enumerate(h) if x.startswith("smsp__average_warps_issue_stalled_")
             and x.endswith("_per_issue_active.ratio")]
    fam = collections.defaultdict(list)
    lines = []
    for r in data:
        name = r[col["Kernel Name"]]
        short = name.split("(")[0].replace("void ", "")
        t = conv(r[col["gpu__time_duration.sum"]], units[col["gpu__time_duration.sum"]])
        dr = conv(r[col["dram__bytes_read.sum"]], units[col["dram__bytes_read.sum"]])
        dw = conv(r[col["dram__bytes_write.sum"]], units[col["dram__bytes_write.sum"]])
        prd = conv(r[col["pcie__read_bytes.sum.per_second"]], units[col["pcie__read_bytes.sum.per_second"]]) * t
        pwr = conv(r[col["pcie__write_bytes.sum.per_second"]], units[col["pcie__write_bytes.sum.per_second"]]) * t
        sysr = conv(r[col["syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum"]], "sector")
        sysw = conv(r[col["syslts__t_sectors_srcunit_tex_aperture_sysmem_op_write_lookup_miss.sum"]], "sector")
        occ = r[col["sm__warps_active.avg.pct_of_peak_sustained_active"]]
        top = sorted(((float(r[i] or 0), h[i][len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")])
                      for i in stall), reverse=True)[:3]
        grid = r[col["launch__grid_size"]]
        lines.append(f"{short:28s} grid={grid:>5s} t={t*1e6:8.2f} us  dram r/w={dr/1e6:7.2f}/{dw/1e6:6.2f} MB  "
                     f"pcie r/w={prd/1e6:6.2f}/{pwr/1e6:6.2f} MB ({prd/t/1e9 if t else 0:5.1f}/{pwr/t/1e9 if t else 0:5.1f} GB/s)  "
                     f"sysmem sectors r/w={sysr/1e6:6.2f}/{sysw/1e6:6.2f} MB  occ={float(occ):5.1f}%  "
                     + " ".join(f"{n}={v:.1f}" for v, n in top))
        fam[short].append(dict(t=t, dram=dr + dw, pcie=prd + pwr, sys=sysr + sysw))
    traffic = {}
    for k, v in fam.items():
        key = k.replace("k_", "").split("<")[0]
        key = {"gather_uniq": "gather", "flush_rows": "urgent", "segreduce": "segred", "dot_model": "model"}.get(key, key)
        host = any(x in k for x in ("gather", "flush"))
        traffic[key] = {"kernel": k, "launches_profiled": len(v),
                        "dram_bytes_per_launch": sum(x["dram"] for x in v) / len(v),
                        "pcie_bytes_per_launch": sum(x["pcie"] for x in v) / len(v),
                        "sysmem_bytes_per_launch": sum(x["sys"] for x in v) / len(v),
                        "traffic_bytes_per_launch": sum(x["dram"] for x in v) / len(v),
                        "traffic_kind": "dram (read+write)",
                        "host_link_bytes_per_launch": sum(x["sys"] for x in v) / len(v) if host else None,
                        "host_link_kind": "sysmem sectors through L2 (read+write)" if host else None}
    open(out_txt, "w").write("\n".join(lines) + "\n")
    json.dump(traffic, open(out_json, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main(*sys.argv[1:4])
