#!/bin/bash
# Fig. 12-shaped ablation on B200 (NEXT-3): the paper's O0 (sample synchronisation, one
# sample per lane), O1 (+ inheritance), O2 (+ warp streaming), against our default
# scheduler (refill threshold 16) with and without streaming.  One JSON line per run.
# usage: bash scripts/ablation.sh > profiles/r01_ablation.jsonl
set -e
cd "$(dirname "$0")/.."
GRID='{"sched": [1, 2, 0], "stream": [0, 1]}'
for cq in "C1 0" "C1 1" "C2 0" "C2 1" "C3 0" "C3 2"; do
    set -- $cq
    python scripts/sweep.py --config "$1" --query "$2" --samples 1e7 --reps 2 --grid "$GRID"
done
