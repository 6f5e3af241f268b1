"""Summarise a gpurun ncu pass into profiles/ (run here, on the CPU box).

    python scripts/summarize_profiles.py r1b
reads  gpurun_out/launches_<tag>.csv   (ncu --metrics gpu__time_duration.sum launch list)
       gpurun_out/prof_<tag>.ncu-rep   (ncu --set full capture of the probe kernels)
       gpurun_out/bench_<tag>.json     (the bench line of the same pass)
writes profiles/<tag>_launches.csv, profiles/<tag>_summary.md, profiles/<tag>_traffic.json
"""
import csv
import io
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("lts__t_requests_srcunit_tex_op_read.sum", "L2 read requests (from SMs)"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from SMs)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("sm__inst_executed.avg.per_cycle_elapsed", "IPC (per SM)"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "long-scoreboard stall / issue"),
]


def launches(tag):
    rows = list(csv.reader(open(os.path.join(OUT, f"launches_{tag}.csv"))))
    i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr = rows[i]
    ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    out = []
    for r in rows[i + 1:]:
        if r[mi] == "gpu__time_duration.sum":
            out.append((int(r[0]), r[ki].split("(")[0].replace("void ", ""),
                        float(r[vi].replace(",", "")) * scale.get(r[ui], 1e-6)))
    return out


def ncu_raw(tag):
    rep = os.path.join(OUT, f"prof_{tag}.ncu-rep")
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    kern = []
    for r in rows[2:]:
        d = {"name": r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "")}
        for m, _ in METRICS:
            if m in hdr:
                d[m] = (r[hdr.index(m)], units[hdr.index(m)])
        kern.append(d)
    return kern


def to_float(v):
    return float(str(v).replace(",", ""))


def main(tag):
    os.makedirs(PROF, exist_ok=True)
    L = launches(tag)
    with open(os.path.join(PROF, f"{tag}_launches.csv"), "w") as f:
        f.write("id,kernel,ms\n")
        for i, n, ms in L:
            if "dyc::" in n:
                f.write(f"{i},{n},{ms:.6f}\n")
    bench = json.load(open(os.path.join(OUT, f"bench_{tag}.json")))
    # the timed steps are the last 2 groups of probe launches before k_gather
    ours = [(n, ms) for _, n, ms in L if "dyc::" in n and "k_gather" not in n and "k_count" not in n]
    starts = [j for j, (n, _) in enumerate(ours) if "k_upsert" in n]
    if any("k_st_scatter<1, 1>" in n for n, _ in ours):
        # a staged insert opens each step: k_st_hist, k_st_scan, k_st_scatter<1, 1>, ...
        starts = [j - 2 for j, (n, _) in enumerate(ours) if "k_st_scatter<1, 1>" in n]
    last2 = ours[starts[-2]:]                      # the last two timed steps
    per = {}
    for n, ms in last2:
        base = n.split("<")[0].replace("dyc::", "")
        per.setdefault(base, []).append(ms)
    step_ms = sum(sum(v) for v in per.values()) / 2
    K = ncu_raw(tag)
    traffic = {}
    md = [f"# Profile summary `{tag}`", "",
          "Source: `gpurun` pass `scripts/gpu_pass.sh " + tag + " ... launches ncu` on one B200 (sm_100a).",
          "",
          "- `ncu --metrics gpu__time_duration.sum --clock-control none`: the launch list of",
          "  `bench.py --steps 2 --warmup 1 --profile-only`. These launches are cold-cache and serialised, so",
          "  compare shares, not absolutes. The full list of our launches is `" + tag + "_launches.csv`.",
          "- `ncu --set full --import-source on -k regex:\"k_upsert|k_find|k_delete|k_place|k_st_\"`: one capture",
          "  per kernel launch of one step (staged passes included), on the same C2 2^27 workload.",
          "", "## Kernel shares of one step (ncu launch list, last two timed steps)", "",
          "| kernel | ms per step | share | bench (CUDA events, warm) ms |", "|---|---|---|---|"]
    kms = bench["roofline"]["kernel_ms_per_step"]
    for base, v in sorted(per.items(), key=lambda x: -sum(x[1])):
        ms = sum(v) / 2
        md.append(f"| {base} | {ms:.3f} | {ms / step_ms:.1%} | {kms.get(base, float('nan')):.3f} |")
    md += ["", "## ncu --set full, per kernel (one launch each)", "",
           "| metric | " + " | ".join(k["name"] for k in K) + " |",
           "|---|" + "---|" * len(K)]
    for m, label in METRICS:
        cells = []
        for k in K:
            v, u = k.get(m, ("", ""))
            cells.append(f"{v} {u}".strip())
        md.append(f"| {label} (`{m}`) | " + " | ".join(cells) + " |")
    for k in K:
        base = k["name"].split("<")[0].replace("dyc::", "")
        try:
            rd = to_float(k["dram__bytes_read.sum"][0]) * (1e9 if k["dram__bytes_read.sum"][1] == "Gbyte" else
                                                          1e6 if k["dram__bytes_read.sum"][1] == "Mbyte" else 1)
            wr = to_float(k["dram__bytes_write.sum"][0]) * (1e9 if k["dram__bytes_write.sum"][1] == "Gbyte" else
                                                           1e6 if k["dram__bytes_write.sum"][1] == "Mbyte" else 1)
            if base not in traffic or rd + wr > traffic[base]:
                traffic[base] = rd + wr
            if base.startswith("k_st_"):       # the bench's profile kind of a staged pass
                kind = {"k_st_hist": "st_hist", "k_st_scan": "st_hist", "k_st_scatter": "st_scatter",
                        "k_st_apply": "st_apply", "k_st_unperm": "st_unperm"}.get(base)
                if kind:
                    traffic[kind] = traffic.get(kind, 0.0) + rd + wr
        except (KeyError, ValueError):
            pass
    r = bench["roofline"]
    md += ["", "## Roofline of the bench line", "",
           f"- Dominant kernel: `{r['kernel']}`, {r['launch_ms']:.3f} ms per launch.",
           f"- Achieved: {r['achieved']:.0f} GB/s of algorithmic bytes.",
           f"  - That is {r['frac']:.3f} of the measured {r['peak']:.0f} GB/s copy peak.",
           f"  - It is {r['frac_of_random_ceiling']:.3f} of the live random-bucket ceiling "
           f"({r['random_bucket_ceiling']['gbs']:.0f} GB/s = {r['random_bucket_ceiling']['gprobes_per_s']:.1f} G bucket reads/s).",
           f"- Traffic (ncu `dram__bytes_read.sum + dram__bytes_write.sum` per launch): "
           f"{traffic.get(r['kernel'], float('nan')) / 1e9:.2f} GB, against "
           f"{r['algorithmic_bytes_per_launch'] / 1e9:.2f} GB algorithmic.",
           "- Per-kernel achieved GB/s (algorithmic bytes ÷ CUDA-event time): "
           + ", ".join(f"{k} {v:.0f}" for k, v in r["achieved_gbs_per_kernel"].items()) + ".",
           ""]
    open(os.path.join(PROF, f"{tag}_summary.md"), "w").write("\n".join(md) + "\n")
    json.dump({k: v for k, v in traffic.items()}, open(os.path.join(PROF, f"{tag}_traffic.json"), "w"), indent=1)
    # the pass bench.py reads its roofline traffic from (tag names do not sort by date)
    json.dump({"tag": tag, "file": f"{tag}_traffic.json"}, open(os.path.join(PROF, "traffic_latest.json"), "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r1")
