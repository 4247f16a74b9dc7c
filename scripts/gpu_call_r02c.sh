#!/bin/bash
# Round-2 measurement call: launch list of the bench command, ncu --set full of both
# sampling kernels at the bench size (and the cyclic query's Alley), the bench line and the
# reference arm.  usage (on the GPU box): bash scripts/gpu_call_r02c.sh r02c
set -u
cd "$(dirname "$0")/.."
TAG=${1:-r02c}
mkdir -p gpurun_out profiles
make all > gpurun_out/${TAG}_build.log 2>&1
bash scripts/profile_round.sh ${TAG} > gpurun_out/${TAG}_profile_round.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:sample_kernel -c 1 \
    -o gpurun_out/${TAG}_cyclic_full python scripts/profile_driver.py --samples 1e7 --query 2 --methods 1 \
    > gpurun_out/${TAG}_cyclic_full.log 2>&1
python scripts/ncu_lines.py gpurun_out/${TAG}_cyclic_full.ncu-rep "" 30 > gpurun_out/${TAG}_cyclic_ncu_lines.txt 2>&1
cp profiles/traffic_latest.json gpurun_out/${TAG}_traffic_latest.json
echo done
