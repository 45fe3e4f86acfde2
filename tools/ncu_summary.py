"""Summarise the ncu outputs brought back by tools/profile_round.sh into profiles/ (committed).

python tools/ncu_summary.py <round tag>   e.g. r01
Writes profiles/<tag>_launches.txt (kernel share of the bench step), profiles/<tag>_ncu_cg.txt
(key counters + stall breakdown of the persistent solve) and profiles/ncu_traffic.json (DRAM bytes
per launch, read by bench.py for the roofline "traffic" field)."""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"


def launches():
    lines = open(os.path.join(OUT, "launches.csv")).read().splitlines()
    i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in csv.DictReader(lines[i:]):
        k = r["Kernel Name"].split("(")[0]
        agg[k][0] += 1
        agg[k][1] += float(r["Metric Value"])
    tot = sum(v[1] for v in agg.values())
    out = ["# ncu --metrics gpu__time_duration.sum --clock-control none, python bench.py --steps 2 --warmup 3",
           "# cold-cache serialised per-launch times: compare SHARES, not absolutes", f"# total {tot/1e6:.3f} ms",
           f"{'ms':>10} {'launches':>8} {'share':>6}  kernel"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{v[1]/1e6:10.3f} {v[0]:8d} {100*v[1]/tot:5.1f}%  {k}")
    return "\n".join(out) + "\n"


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(txt)))
    return {h: (u, v) for h, u, v in zip(r[0], r[1], r[2])}


def to_bytes(u, v):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)


def stalls(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(txt)))
    h, rows = r[1], r[2:]
    names = [n for n in h if n.startswith("stall_") and "Not Issued" not in n]
    tot = {n: sum(int(x[h.index(n)] or 0) for x in rows) for n in names}
    T = sum(tot.values()) or 1
    return ", ".join(f"{n[6:]} {100*v/T:.1f}%" for n, v in sorted(tot.items(), key=lambda x: -x[1])[:8])


def main():
    os.makedirs(PROF, exist_ok=True)
    if os.path.exists(os.path.join(OUT, "launches.csv")):
        open(os.path.join(PROF, f"{tag}_launches.txt"), "w").write(launches())
    rep = os.path.join(OUT, "prof_cg_dyn.ncu-rep")
    if os.path.exists(rep):
        m = raw(rep)
        keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
                "l1tex__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
                "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
                "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
                "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum",
                "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
        lines = ["# ncu --set full --clock-control none: cg_persistent<DYN> (whole C2 solve, one launch),",
                 "# python tools/one_solve.py C2 1 2 (dynamic mixed precision)"]
        for k in keys:
            if k in m:
                lines.append(f"{k:60s} {m[k][1]:>20s} {m[k][0]}")
        lines.append("stall breakdown (all samples): " + stalls(rep))
        open(os.path.join(PROF, f"{tag}_ncu_cg.txt"), "w").write("\n".join(lines) + "\n")
        dram = to_bytes(*m["dram__bytes_read.sum"]) + to_bytes(*m["dram__bytes_write.sum"])
        tp = os.path.join(PROF, "ncu_traffic.json")
        d = json.load(open(tp)) if os.path.exists(tp) else {}
        d["C2"] = {"dram_bytes_per_launch": dram, "kernel": "cg_persistent<DYN> (one launch = one whole solve)",
                   "source": f"profiles/{tag}_ncu_cg.txt"}
        json.dump(d, open(tp, "w"), indent=1)
        print("\n".join(lines))
    # DRAM traffic of the other configs' persistent solves (tools/gpu_final_r2.sh: ncu --metrics
    # dram__bytes_read.sum,dram__bytes_write.sum on one solve each, gpurun_out/traffic_<cfg>.csv)
    tp = os.path.join(PROF, "ncu_traffic.json")
    d = json.load(open(tp)) if os.path.exists(tp) else {}
    for f in sorted(os.listdir(OUT)):
        if not (f.startswith("traffic_") and f.endswith(".csv")):
            continue
        cfg = f[len("traffic_"):-4]
        lines = open(os.path.join(OUT, f)).read().splitlines()
        hdr = [k for k, l in enumerate(lines) if l.startswith('"ID"')]
        if not hdr:
            continue
        tot, kern = 0.0, None
        for r in csv.DictReader(lines[hdr[0]:]):
            if "_persistent" not in r["Kernel Name"]:
                continue
            kern = r["Kernel Name"].split("(")[0]
            tot += to_bytes(r["Metric Unit"], r["Metric Value"])
        if kern:
            d[cfg] = {"dram_bytes_per_launch": tot, "kernel": kern + " (one launch = one whole solve)",
                      "source": f"profiles/{tag}_traffic_{cfg}.csv"}
            open(os.path.join(PROF, f"{tag}_traffic_{cfg}.csv"), "w").write("\n".join(lines[hdr[0]:]) + "\n")
            print(cfg, kern, f"{tot/1e9:.3f} GB per launch")
    json.dump(d, open(tp, "w"), indent=1)


if __name__ == "__main__":
    main()
