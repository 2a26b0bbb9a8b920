#!/bin/bash
# compute-sanitizer over the C1-sized GPU parity tests (sampling, graph-replayed steps, replicated and tiered
# gathers, bucketing, logical-rank relay): memcheck, racecheck, synccheck, initcheck. (No leak check: the
# torch caching allocator keeps its segments until process exit by design.)
# Usage: bash tools/sanitize.sh [outdir]   -> one log per tool + a summary line each
OUT=${1:-gpurun_out/sanitize}
mkdir -p "$OUT"
SEL="step_batch or bind_step or one_local_bin_with_placement or c1_full_size or handmade or empty_batch or tiered_and_bucket or group_relay or step_graph or step_host or gather_replicated or reused_ctx or replicated_hot or sage_mean_on_sampled"
# initcheck shadows every byte torch allocates (slow): it runs on the hand-made graphs and an empty batch only
for tool in memcheck racecheck synccheck initcheck; do
    sel="$SEL"
    [ "$tool" = initcheck ] && sel="handmade or empty_batch"
    timeout 1200 compute-sanitizer --tool $tool --target-processes all --print-limit 50 \
        python -m pytest tests/test_gpu_parity.py tests/test_gpu_sage.py -x -q -k "$sel" -p no:cacheprovider > "$OUT/$tool.log" 2>&1
    echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' "$OUT/$tool.log" | sort | uniq -c | tr '\n' ' ') $(grep -E 'passed|failed' "$OUT/$tool.log" | tail -1)"
done | tee "$OUT/summary.txt"
