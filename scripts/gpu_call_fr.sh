#!/bin/bash
# GPU call: frontier parity tests + A/B timing
set -u
cd "$(dirname "$0")/.."
TAG=${1:-fr}
mkdir -p gpurun_out
make all > gpurun_out/${TAG}_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_frontier.py -q -x -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
timeout 1200 python scripts/frontier_ab.py ${AB_ARGS:-} > gpurun_out/${TAG}_ab.jsonl 2> gpurun_out/${TAG}_ab.err
echo "ab rc=$?" >> gpurun_out/${TAG}_ab.err
echo done
