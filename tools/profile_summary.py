"""Summarise an ncu capture and launch list into profiles/ (committed evidence for the bench roofline).

    python tools/profile_summary.py TAG            # reads gpurun_out/prof_TAG.ncu-rep, launches_TAG.csv
        -> profiles/TAG_ncu_summary.json, profiles/TAG_ncu_full_summary.txt, profiles/TAG_launches.csv

The launch list is `ncu --metrics gpu__time_duration.sum --clock-control none` of a short bench run
(cold-cache, serialised launches: compare the SHARE of each kernel, not absolute times).  The full capture
gives per-kernel DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum), the `traffic` of the roofline.
"""
import collections
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1.0, "ms": 1e3}
WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "smsp__inst_executed.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]


def short(name):
    for k in ("vpps_df", "vpps_cl", "vpps_fb", "vpps_dw_gemm", "vpps_leaf_fwd", "sgd_kernel", "FillFunctor"):
        if k in name:
            return k
    return name[:40]


def main():
    tag = sys.argv[1]
    out_dir = os.path.join(ROOT, "profiles")
    rep = os.path.join(ROOT, "gpurun_out", f"prof_{tag}.ncu-rep")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    head, units = rows[0], rows[1]
    kernels = collections.OrderedDict()
    for r in rows[2:]:
        name = short(r[head.index("Kernel Name")])
        d = {}
        for w in WANT:
            if w in head:
                i = head.index(w)
                try:
                    v = float(r[i])
                except ValueError:
                    continue
                u = units[i]
                if u in SCALE and ("bytes" in w or "duration" in w):
                    v *= SCALE[u]
                d[w] = v
        kernels.setdefault(name, []).append(d)
    summary = {"tag": tag, "capture": "ncu --set full --clock-control none (caches flushed per replay)",
               "kernels": {}}
    for k, lst in kernels.items():
        avg = {w: sum(x.get(w, 0.0) for x in lst) / len(lst) for w in WANT if any(w in x for x in lst)}
        avg["dram_bytes_per_launch"] = avg.get("dram__bytes_read.sum", 0.0) + avg.get("dram__bytes_write.sum", 0.0)
        avg["launches_captured"] = len(lst)
        summary["kernels"][k] = avg
    dom = "vpps_df" if "vpps_df" in summary["kernels"] else next(iter(summary["kernels"]))
    summary["dominant_kernel"] = dom
    summary["dram_bytes_per_launch"] = summary["kernels"][dom]["dram_bytes_per_launch"]
    launches = os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv")
    if os.path.exists(launches):
        lrows = [r for r in csv.DictReader(l for l in open(launches) if not l.startswith("=="))]
        per = collections.defaultdict(list)
        for r in lrows:
            if r.get("Metric Name") == "gpu__time_duration.sum":
                v = float(r["Metric Value"]) * SCALE.get(r.get("Metric Unit", "ns"), 1e-3)
                per[short(r["Kernel Name"])].append(v)
        tot = sum(sum(v) for k, v in per.items() if k != "FillFunctor")
        summary["launch_list_us"] = {k: {"n": len(v), "mean_us": sum(v) / len(v),
                                         "share_of_step": (sum(v) / tot if k != "FillFunctor" else None)}
                                     for k, v in per.items()}
        shutil.copy(launches, os.path.join(out_dir, f"{tag}_launches.csv"))
    # in-pipeline DRAM (ncu --cache-control none over a bench run, L2 flush kernel between steps): what a
    # real pass reads from / writes to DRAM; writes include evictions of the flush buffer's dirty lines
    inpipe = os.path.join(ROOT, "gpurun_out", f"dram_inpipe_{tag}.csv")
    if os.path.exists(inpipe):
        lrows = [r for r in csv.DictReader(l for l in open(inpipe) if not l.startswith("=="))]
        per = collections.defaultdict(lambda: collections.defaultdict(list))
        for r in lrows:
            v = float(r["Metric Value"]) * SCALE.get(r.get("Metric Unit", "byte"), 1.0)
            per[short(r["Kernel Name"])][r["Metric Name"]].append(v)
        ip = {k: {m: sum(l) / len(l) for m, l in d.items()} | {"launches": len(next(iter(d.values())))}
              for k, d in per.items()}
        pass_k = [k for k in ip if k != "FillFunctor"]
        summary["in_pipeline"] = {
            "capture": "ncu --cache-control none --clock-control none (bench steps, 256 MiB L2 flush between steps)",
            "kernels": ip,
            "pass_dram_read_bytes": sum(ip[k].get("dram__bytes_read.sum", 0.0) for k in pass_k),
            "pass_dram_write_bytes": sum(ip[k].get("dram__bytes_write.sum", 0.0) for k in pass_k)}
        shutil.copy(inpipe, os.path.join(out_dir, f"{tag}_dram_inpipe.csv"))
    with open(os.path.join(out_dir, f"{tag}_ncu_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
    details = subprocess.run(["ncu", "-i", rep, "--page", "details"], capture_output=True, text=True).stdout
    with open(os.path.join(out_dir, f"{tag}_ncu_full_summary.txt"), "w") as f:
        f.write(details)
    print(json.dumps({k: {"us": v.get("gpu__time_duration.sum"), "dram_MB": v["dram_bytes_per_launch"] / 1e6}
                      for k, v in summary["kernels"].items()}, indent=1))


if __name__ == "__main__":
    main()
