#!/bin/bash
set -u
cd "$(dirname "$0")/.."
TAG=${1:-frp}
mkdir -p gpurun_out
make all > gpurun_out/${TAG}_build.log 2>&1
for Q in 1 0; do
timeout 600 ncu --metrics gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread,launch__occupancy_limit_registers --clock-control none --profile-from-start off --csv \
   --log-file gpurun_out/${TAG}_q${Q}_levels.csv python scripts/profile_driver.py --samples 4194304 --path 1 --query $Q --methods 1 > gpurun_out/${TAG}_q${Q}_levels.log 2>&1
done
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:frontier_kernel -c 7 \
    -o gpurun_out/${TAG}_full python scripts/profile_driver.py --samples 4194304 --path 1 --query 1 --methods 1 > gpurun_out/${TAG}_full.log 2>&1
python scripts/ncu_lines.py gpurun_out/${TAG}_full.ncu-rep "" 25 > gpurun_out/${TAG}_lines.txt 2>&1
echo done
