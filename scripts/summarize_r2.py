"""Turns the bench lines of `scripts/gpu_pass.sh TAG ablation sweeps` into the
markdown tables of profiles/r2_ablation.md and profiles/r2_sweeps.md.

    python scripts/summarize_r2.py TAG
"""
import glob
import json
import os
import sys

OUT = "gpurun_out"


def load(path):
    try:
        lines = [l for l in open(path).read().splitlines() if l.startswith("{")]
        return json.loads(lines[-1]) if lines else None
    except OSError:
        return None


def c2_row(x):
    t = x["table"]
    ops = x["ops"]
    return (f"{x['value']:,.0f} | {ops['insert_mops']:,.0f} | {ops['find_mops']:,.0f} | {ops['delete_mops']:,.0f} | "
            f"{t['phi']:.3f} | {t['evictions_per_insert']:.3f} | "
            f"{'/'.join(f'{f:.2f}' for f in t['per_table_fill'])}")


def ablation(tag):
    rows = ["| placement | d | B | step Mops/s | insert | find | delete | φ | evictions per insert | per-table fill |",
            "|---|---|---|---|---|---|---|---|---|---|"]
    for pl in ("first_fit", "paper_weighted"):
        for suffix, d, B in [(f"d{d}", d, 8) for d in (2, 3, 4, 6, 8)] + [("B4", 4, 4), ("B16", 4, 16)]:
            x = load(os.path.join(OUT, f"abl_{tag}_{pl}_{suffix}.json"))
            if x:
                rows.append(f"| {pl} | {d} | {B} | {c2_row(x)} |")
    rows += ["", "C3-RE (x0.25), whole stream:", "",
             "| placement | Mops/s | insert | find | delete | φ at peak | per-table fill at peak | evictions per new key | host waits / batch |",
             "|---|---|---|---|---|---|---|---|---|"]
    for pl in ("first_fit", "paper_weighted"):
        x = load(os.path.join(OUT, f"abl_{tag}_{pl}_c3.json"))
        if x:
            o, p = x["ops"], x["at_peak_live"]
            rows.append(f"| {pl} | {x['value']:,.0f} | {o.get('insert_mops', 0):,.0f} | {o.get('find_mops', 0):,.0f} | "
                        f"{o.get('delete_mops', 0):,.0f} | {p['phi']:.3f} | "
                        f"{'/'.join(f'{f:.2f}' for f in p['per_table_fill'])} | "
                        f"{p['evictions_per_new_key_whole_stream']:.3f} | {x.get('host_waits_per_batch')} |")
    return "\n".join(rows)


def sweeps(tag):
    rows = ["| θ | step Mops/s | insert | find | delete | φ | evictions per insert | per-table fill |",
            "|---|---|---|---|---|---|---|---|"]
    for th in ("0.7", "0.75", "0.8", "0.85", "0.9"):
        x = load(os.path.join(OUT, f"sw_{tag}_theta{th}.json"))
        if x:
            rows.append(f"| {th} | {c2_row(x)} |")
    rows += ["", "| parameter | Mops/s | insert | find | delete | min fill after a mutation | max fill | peak table MB | host waits / batch |",
             "|---|---|---|---|---|---|---|---|---|"]
    for f in sorted(glob.glob(os.path.join(OUT, f"sw_{tag}_c3*.json"))):
        x = load(f)
        if not x:
            continue
        name = os.path.basename(f)[len(f"sw_{tag}_c3"):-5].strip("_").replace("_", " ")
        o, ft = x["ops"], x["fill_track"]
        rows.append(f"| {name} | {x['value']:,.0f} | {o.get('insert_mops', 0):,.0f} | {o.get('find_mops', 0):,.0f} | "
                    f"{o.get('delete_mops', 0):,.0f} | {ft['min_after_mutation']:.3f} | {ft['max']:.3f} | "
                    f"{x['table_bytes']['max'] / 2**20:.1f} | {x.get('host_waits_per_batch')} |")
    return "\n".join(rows)


if __name__ == "__main__":
    tag = sys.argv[1]
    print("## Ablation\n")
    print(ablation(tag))
    print("\n## Sweeps\n")
    print(sweeps(tag))
