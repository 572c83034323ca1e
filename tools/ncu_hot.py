"""Summarise an ncu report: key raw metrics, stall reasons and the hottest SASS lines.
usage: python tools/ncu_hot.py gpurun_out/prof_TAG.ncu-rep [n_top]"""
import collections, csv, io, subprocess, sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 30
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__registers_per_thread",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum", "smsp__cycles_active.avg",
        "sm__cycles_elapsed.avg"]
for i, h in enumerate(hdr):
    if h in keys:
        print(f"{h:60s} {vals[i]:>16s} {units[i]}")
st = {h: float(vals[i]) for i, h in enumerate(hdr) if h.startswith("smsp__pcsamp_warps_issue_stalled_")
      and not h.endswith("not_issued") and vals[i] not in ("", "n/a")}
tot = sum(st.values()) or 1
print("stalls:", ", ".join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_','')} {v/tot*100:.1f}%"
                           for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:10]))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(src)))
h = r[1]
d = r[2:]
ia, isrc, isamp, iex = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), \
    h.index("Instructions Executed")
tot = sum(float(x[isamp] or 0) for x in d)
for x in sorted(d, key=lambda x: -float(x[isamp] or 0))[:ntop]:
    print(f"{x[ia][-5:]} {float(x[isamp])/tot*100:5.1f}% {x[iex]:>9s} {x[isrc][:80]}")
c = collections.Counter()
for x in d:
    op = [o for o in x[isrc].split() if not o.startswith("@")]
    c[op[0].split(".")[0] if op else ""] += float(x[iex] or 0)
t = sum(c.values())
print("instr mix:", ", ".join(f"{k} {v/t*100:.1f}%" for k, v in c.most_common(12)), f"total {t/1e6:.1f}M")
