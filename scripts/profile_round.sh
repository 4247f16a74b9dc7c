#!/bin/bash
# One GPU call that refreshes every committed measurement of the bench workload:
#   1. ncu launch list of the bench command (cold-cache, serialised: compare shares);
#   2. ncu --set full of both sampling kernels at the bench size (1e8 samples), with
#      source correlation, summarised into profiles/<tag>_ncu_details.json and
#      profiles/traffic_latest.json (DRAM bytes per sample -> the bench's "traffic");
#   3. the bench line itself (never under a profiler).
# usage (on the GPU box): bash scripts/profile_round.sh r01b
set -u
cd "$(dirname "$0")/.."
TAG=${1:-latest}
mkdir -p gpurun_out profiles
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-qerror --no-cyclic \
    > gpurun_out/${TAG}_launches_bench.log 2>&1
# profile_driver brackets the two bench-size launches with cudaProfilerStart/Stop
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:sample_kernel -c 2 \
    -o gpurun_out/${TAG}_full python scripts/profile_driver.py --samples 1e8 > gpurun_out/${TAG}_full.log 2>&1
python scripts/ncu_summary.py gpurun_out/${TAG}_full.ncu-rep profiles/${TAG}_ncu_details.json 1e8 \
    > gpurun_out/${TAG}_summary.log 2>&1
python scripts/launch_summary.py gpurun_out/${TAG}_launches.csv > gpurun_out/${TAG}_launches_summary.md 2>&1
python scripts/ncu_lines.py gpurun_out/${TAG}_full.ncu-rep "" 30 > gpurun_out/${TAG}_ncu_lines.txt 2>&1
cp profiles/${TAG}_ncu_details.json profiles/traffic_latest.json gpurun_out/ 2>/dev/null
timeout 900 python bench.py > gpurun_out/${TAG}_bench.jsonl 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference > gpurun_out/${TAG}_bench_reference.jsonl 2> gpurun_out/${TAG}_bench_reference.err
echo done
