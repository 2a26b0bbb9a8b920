"""Markdown table of tools/sim_plan.py's predictions.
    python tools/sim_table.py [profiles/r01_plan_sim.jsonl] [--switch 1]
"""
import json
import sys


def main():
    path = next((a for a in sys.argv[1:] if not a.startswith("--")), "profiles/r01_plan_sim.jsonl")
    gps = int(sys.argv[sys.argv.index("--switch") + 1]) if "--switch" in sys.argv else 1
    print("| Config | k | DDAK: T* us (ingest / NVLink / HBM) | + replicas: best r, T* us (ingest / NVLink / HBM) "
          "| predicted M seeds/s DDAK -> best |")
    print("|---|---|---|---|---|")
    last = None
    for line in open(path):
        d = json.loads(line)
        if d["gpus_per_switch"] != gps:
            continue
        b, bb = d["ddak"], d["ddak_replicated"]
        name = d["config"] if d["config"] != last else ""
        last = d["config"]
        r = d["best_r"]
        rs = "0" if r == 0 else (f"{r / 1e6:.2f} M" if r >= 1e5 else str(r))
        p0, p1 = d["pred_seeds_per_s_ddak"] / 1e6, d["pred_seeds_per_s_best"] / 1e6
        pred = f"{p0:.3g}" if abs(p0 - p1) < 1e-9 else f"{p0:.3g} -> {p1:.3g}"
        print(f"| {name} | {d['k']} | {b['t_star']} ({b['t_ingest']} / {b['t_nvlink']} / {b['t_hbm']}) | "
              f"{rs}, {bb['t_star']} ({bb['t_ingest']} / {bb['t_nvlink']} / {bb['t_hbm']}) | {pred} |")


if __name__ == "__main__":
    main()
