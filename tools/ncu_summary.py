"""Summarise `ncu --set full` reports of one bench config (exported with
`ncu -i X.ncu-rep --page raw --csv --print-units base`, so every value is in base units:
bytes, ns, bytes/s, sectors): per kernel launch the duration, DRAM bytes, PCIe bytes (rate x
duration), sysmem sectors, occupancy and the top stall reasons.  Each figure is checked
against its physical ceiling (DRAM <= 1.1 x the measured HBM peak, PCIe <= 70 GB/s per
direction) and the run fails loudly otherwise -- round 1 mis-scaled auto-unit CSVs.

Updates profiles/ncu_traffic.json[config] = {source_sha, file, kernels: {phase: per-launch
means}}; bench.py reports roofline.traffic from it only while source_sha matches the
benched source.

    python tools/ncu_summary.py CONFIG OUT_TXT RAW_CSV [RAW_CSV ...]
"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
PHASE = {"k_gather_uniq": "gather", "k_flush_rows": "urgent", "k_segreduce": "segred", "k_dot_model": "model",
         "k_update1": "segred", "k_dot_rg": "model", "k_pack_drain": "side",
         "k_expand": "expand", "k_segred_combine": "segred_combine", "k_segred_chunks": "segred_chunks",
         "k_schedule": "schedule", "k_optimizer": "optimizer", "k_transe_pos": "model_pos",
         "k_transe_pairs_tiled": "model_pairs", "k_transe_grads_tiled": "model_grads"}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {"hbm_gbs": 6554.6}


def read_rows(path):
    rows = list(csv.reader(open(path)))
    h = rows[0]
    units = rows[1]
    data = [r for r in rows[2:] if len(r) == len(h)]
    return h, units, data


def main(config, out_txt, *raws):
    hbm = peaks()["hbm_gbs"] * 1e9
    fam = collections.defaultdict(list)
    lines, bad = [], []
    for raw in raws:
        h, units, data = read_rows(raw)
        col = {n: i for i, n in enumerate(h)}
        if "gpu__time_duration.sum" not in col:  # no launch matched (e.g. k_expand with the fused lookup)
            print(f"# {raw}: no report, skipped")
            continue
        for need, unit in [("gpu__time_duration.sum", "ns"), ("dram__bytes_read.sum", "byte"),
                           ("dram__bytes_write.sum", "byte")]:
            u = units[col[need]]
            if u != unit:
                sys.exit(f"{raw}: {need} is in '{u}', not base unit '{unit}': export with --print-units base")
        stall = [i for i, x in enumerate(h) if x.startswith("smsp__average_warps_issue_stalled_")
                 and x.endswith("_per_issue_active.ratio")]
        f = lambda r, n: float(r[col[n]].replace(",", "") or 0) if n in col else 0.0
        for r in data:
            name = r[col["Kernel Name"]]
            short = name.split("(")[0].replace("void ", "").replace("frugal::", "")
            t = f(r, "gpu__time_duration.sum") * 1e-9
            dr, dw = f(r, "dram__bytes_read.sum"), f(r, "dram__bytes_write.sum")
            prd = f(r, "pcie__read_bytes.sum.per_second") * t
            pwr = f(r, "pcie__write_bytes.sum.per_second") * t
            sysr = f(r, "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum") * 32
            sysw = f(r, "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_write_lookup_miss.sum") * 32
            occ = f(r, "sm__warps_active.avg.pct_of_peak_sustained_active")
            top = sorted(((float(r[i] or 0), h[i][len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")])
                          for i in stall), reverse=True)[:3]
            grid = r[col["launch__grid_size"]]
            line = (f"{short:34s} grid={grid:>5s} t={t*1e6:8.2f} us  dram r/w={dr/1e6:7.2f}/{dw/1e6:6.2f} MB "
                    f"({(dr+dw)/t/1e9 if t else 0:6.0f} GB/s)  pcie r/w={prd/1e6:6.2f}/{pwr/1e6:6.2f} MB "
                    f"({prd/t/1e9 if t else 0:5.1f}/{pwr/t/1e9 if t else 0:5.1f} GB/s)  sysmem r/w={sysr/1e6:6.2f}/"
                    f"{sysw/1e6:6.2f} MB  occ={occ:5.1f}%  " + " ".join(f"{n}={v:.1f}" for v, n in top))
            if t and ((dr + dw) / t > 1.1 * hbm or prd / t > 70e9 or pwr / t > 70e9):
                bad.append(line)
            lines.append(line)
            fam[short.split("<")[0]].append(dict(kernel=short, t=t, dram=dr + dw, pcie=prd + pwr, sys=sysr + sysw))
    if bad:
        sys.exit("figures above their physical ceiling (unit error?):\n" + "\n".join(bad))
    kernels = {}
    for k, v in fam.items():
        key = PHASE.get(k, k)
        host = any(x in k for x in ("gather", "flush"))
        n = len(v)
        kernels[key] = {"kernel": v[0]["kernel"], "launches_profiled": n,
                        "time_us_per_launch": sum(x["t"] for x in v) / n * 1e6,
                        "dram_bytes_per_launch": sum(x["dram"] for x in v) / n,
                        "pcie_bytes_per_launch": sum(x["pcie"] for x in v) / n,
                        "sysmem_bytes_per_launch": sum(x["sys"] for x in v) / n,
                        "traffic_bytes_per_launch": sum(x["dram"] for x in v) / n,
                        "traffic_kind": "dram (read+write)",
                        "host_link_bytes_per_launch": sum(x["sys"] for x in v) / n if host else None,
                        "host_link_kind": "sysmem sectors through L2 (read+write)" if host else None}
    import bench
    jp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        allj = json.load(open(jp))
        if "kernels" not in next(iter(allj.values()), {}):
            allj = {}  # round-1 flat format: superseded
    except Exception:
        allj = {}
    allj[config] = {"source_sha": bench.source_sha(), "file": os.path.relpath(out_txt, ROOT), "kernels": kernels}
    json.dump(allj, open(jp, "w"), indent=1)
    open(out_txt, "w").write(f"# config {config}, source sha {bench.source_sha()}, base units\n" + "\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main(*sys.argv[1:])
