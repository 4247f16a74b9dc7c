#!/bin/bash
# One GPU call: GPU test suite, smoke, bench line (never under a profiler).
# usage (on the GPU box): bash scripts/gpu_call_r02.sh r02a
set -u
cd "$(dirname "$0")/.."
TAG=${1:-r02}
mkdir -p gpurun_out
make all > gpurun_out/${TAG}_build.log 2>&1
timeout 2700 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 1200 python bench.py > gpurun_out/${TAG}_bench.jsonl 2> gpurun_out/${TAG}_bench.err
echo "bench rc=$?" >> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference > gpurun_out/${TAG}_bench_reference.jsonl 2> gpurun_out/${TAG}_bench_reference.err
echo done
