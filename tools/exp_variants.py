"""Runtime variants of the step on ONE resident State (graph + table built once): for each setting of
MOMENT_* environment knobs read at ctx creation, the lanes are re-created and the sampling-only and full step
us per batch measured (tools/sampler_roofline.py's loop), interleaved `--reps` times.

    python tools/exp_variants.py --config C3 --lanes 8 MOMENT_COMPACT_MODE=0 MOMENT_COMPACT_MODE=1 ...
    (a setting may hold several knobs joined by commas: A=1,B=2; "-" = no knob)
"""
import argparse
import gc
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
sys.path.insert(0, os.path.join(ROOT, "tools"))
import sampler_roofline as SR  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--lanes", type=int, default=16)
    ap.add_argument("--batches", type=int, default=2000)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("settings", nargs="+")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, a.lanes)
    streams = [L.stream for L in st.lanes]
    dev = st.device
    out = []
    for rep in range(a.reps):
        for setting in a.settings:
            kv = [] if setting == "-" else [x.split("=", 1) for x in setting.split(",")]
            saved = {k: os.environ.get(k) for k, _ in kv}
            os.environ.update({k: v for k, v in kv})
            st.lanes = None
            gc.collect()
            torch.cuda.empty_cache()
            st.lanes = [bench.Lane(st.M, st.cfg, st.fanout, st.B, st.R, 0, 1, dev, st.table, s) for s in streams]
            for k, v in saved.items():
                if v is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = v
            us_s = SR.timed(st, a.batches, False)
            us_f = SR.timed(st, a.batches, True)
            r = {"setting": setting, "rep": rep, "sampling_only_us": round(us_s, 2), "full_step_us": round(us_f, 2),
                 "seeds_per_s_M": round(st.B / us_f, 3)}
            out.append(r)
            print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
